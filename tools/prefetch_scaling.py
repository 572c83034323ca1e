"""Host script-builder throughput with 1-4 prefetch workers (plan-only model, TGT batches)."""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_micro_khorasanieas18_b200 import vpps  # noqa: E402

print("cpus:", os.cpu_count(), "affinity:", len(os.sched_getaffinity(0)))
m = vpps.Model("binary", 256, 256, 5, n_sm=144, groups=9, plan_only=True, cluster=16, dataflow=True)
csr = [vpps.CsrBatch.from_graphs(synth.config_batch("tgt", i)) for i in range(64)]
for w in (1, 2, 3, 4, 6):
    t = time.perf_counter()
    n = sum(1 for _ in vpps.prefetch_scripts(m, (csr[k % 64] for k in range(400)), workers=w))
    print(f"workers {w}: {(time.perf_counter() - t) / n * 1e6:.1f} us/script")
