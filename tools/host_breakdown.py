"""Fig.10-style CPU/GPU breakdown: the script builder's phases on one host
core for the bench's 64 TGT batches (tools/host_breakdown.cpp, script.cpp built with -DVPPS_HOST_PHASES),
next to the device step time of the bench.
    python tools/host_breakdown.py [bench.json]"""
import json
import os
import subprocess
import sys
import tempfile

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_micro_khorasanieas18_b200 import vpps  # noqa: E402

tmp = tempfile.mkdtemp()
data = os.path.join(tmp, "batches.bin")
with open(data, "wb") as f:
    f.write(np.int32(64).tobytes())
    for b in range(64):
        for a in vpps.CsrBatch.from_graphs(synth.config_batch("tgt", b)).arrays:
            a = np.ascontiguousarray(a, dtype=np.int32)
            f.write(np.int32(len(a)).tobytes())
            f.write(a.tobytes())
exe = os.path.join(tmp, "host_breakdown")
host = os.path.join(ROOT, "paper_conf_micro_khorasanieas18_b200", "csrc", "host")
subprocess.run(["g++", "-O3", "-std=c++17", "-DVPPS_HOST_PHASES", "-I", host, os.path.join(ROOT, "tools", "host_breakdown.cpp"),
                os.path.join(host, "script.cpp"), "-o", exe], check=True)
out = subprocess.run([exe, data, "20"], capture_output=True, text=True, check=True).stdout
print(out, end="")
if len(sys.argv) > 1:
    d = json.load(open(sys.argv[1]))
    print(f"device step (bench, kernels only)        {1e3 * d['ms_per_step']:8.1f} us; e2e step {16e6 / d['e2e']['value']:.1f} us "
          f"with 3 builder threads")
