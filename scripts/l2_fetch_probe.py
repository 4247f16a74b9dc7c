"""L2 fetch-granularity probe: cudaLimitMaxL2FetchGranularity (a hint, 0..128 bytes) set in the
process before the context is created, then the K5 random-gather rates and the C1 sampling
kernels.  One child process per setting.  usage: python scripts/l2_fetch_probe.py [32 64 128 -1]"""
import json
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import json, os, sys
sys.path.insert(0, %r)
import torch
from cuda.bindings import runtime as rt
gran = int(os.environ["GRAN"])
torch.cuda.init(); torch.empty(1, device="cuda")
if gran >= 0:
    err, = rt.cudaDeviceSetLimit(rt.cudaLimit.cudaLimitMaxL2FetchGranularity, gran)
err, cur = rt.cudaDeviceGetLimit(rt.cudaLimit.cudaLimitMaxL2FetchGranularity)
import paper_journals_pacmmod_yelsg24_b200 as G
from workloads import gen
out = {"set": gran, "limit": int(cur)}
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
with G.Context(0) as ctx:
    out["gather"] = {mb: ctx.gather_roofline(mb << 20, 4) for mb in (64, 128, 450, 2048)}
    g, qs = gen.CONFIGS["C1"]()
    ctx.load_graph_obj(g)
    for qi in (1, 2):
        ctx.load_query_obj(qs[qi])
        for m in (G.WJ, G.ALLEY):
            ctx.estimate(m, 2_000_000, 1)
            ts = []
            for rep in range(3):
                flush.fill_(rep); torch.cuda.synchronize()
                r = ctx.estimate(m, 100_000_000, 42)
                ts.append(ctx.last_kernel_seconds())
            out[f"q{qi}_m{m}_ms"] = 1e3 * min(ts)
            out[f"q{qi}_m{m}_est"] = r["estimate"]
print(json.dumps(out), flush=True)
""" % HERE

for gran in (sys.argv[1:] or ["-1", "32", "64", "128"]):
    subprocess.run([sys.executable, "-c", CHILD], env=dict(os.environ, GRAN=gran), check=False)
