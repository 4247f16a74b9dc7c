"""A/B timing of compile-time kernel variants (`make variant OUT=... XFLAGS=-D...`):
each library runs in its own process (GSWORD_LIB) on the same workloads; one JSON line
per (library, workload, query, method) with the best-of-reps sampling-kernel time.
usage: python scripts/variant_bench.py build/variants/lib_a.so build/variants/lib_b.so"""
import json
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r"""
import json, os, sys
sys.path.insert(0, %r)
import torch
import paper_journals_pacmmod_yelsg24_b200 as G
from workloads import gen
N = int(float(os.environ.get("VB_SAMPLES", "1e8")))
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
work = [w.split(":") for w in os.environ.get("VB_WORK", "C1:1,C1:0,C2:0").split(",")]
cache = {}
with G.Context(0) as ctx:
    opts = [o.split("=") for o in os.environ.get("VB_OPTS", "").split(",") if o]
    for k, v in opts:  # gsword_set_option(id, value) before any load, e.g. VB_OPTS=11=32
        ctx.set_option(int(k), int(v))
    for cfg, qi in work:
        if cfg not in cache:
            cache[cfg] = gen.CONFIGS[cfg]()
        g, qs = cache[cfg]
        ctx.load_graph_obj(g)
        ctx.load_query_obj(qs[int(qi)])
        for m in (G.WJ, G.ALLEY):
            ctx.estimate(m, 2_000_000, 1)
            ts = []
            for rep in range(3):
                flush.fill_(rep)
                torch.cuda.synchronize()
                r = ctx.estimate(m, N, 42)
                ts.append(ctx.last_kernel_seconds())
            print(json.dumps({"lib": os.path.basename(G.gsword.LIB_PATH) + os.environ.get("VB_TAG", ""), "config": cfg, "query": int(qi), "method": m,
                              "kernel_ms": 1e3 * min(ts), "samples_per_s": N / min(ts), "est": r["estimate"],
                              "valid": r["n_valid"], "tuned": ctx.query_info()}), flush=True)
""" % HERE

for lib in sys.argv[1:]:
    env = dict(os.environ, GSWORD_LIB=os.path.abspath(lib))
    subprocess.run([sys.executable, "-c", CHILD], env=env, check=False)
