"""Create one handle on a GPU-generated workload and run it R times (builder tooling for ncu).

usage: python scripts/prof_run.py [--workload rmat] [--scale 26] [--runs 1] [--round-loop 0]
"""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import graphgen.gpu as gg
import paper_conf_sc_mandulakgfhs24_b200 as lm

p = argparse.ArgumentParser()
p.add_argument("--workload", default="rmat")
p.add_argument("--scale", type=int, default=26)
p.add_argument("--runs", type=int, default=1)
p.add_argument("--round-loop", type=int, default=0)
p.add_argument("--key-cache", action="store_true")
a = p.parse_args()
dev = torch.device("cuda:0")
torch.cuda.set_device(dev)
if a.workload == "rmat":
    dg = gg.rmat(a.scale, 16, seed=1, weights="uniform", device=dev)
elif a.workload == "er":
    dg = gg.er(1 << a.scale, 16.0, seed=1, weights="uniform", device=dev)
else:
    side = 1 << (a.scale // 2)
    dg = gg.mesh(side, keep=0.6 if a.workload == "road" else 1.0, seed=1,
                 weights="gradient" if a.workload == "gradient" else "uniform", device=dev)
stream = torch.cuda.current_stream(dev).cuda_stream
opts = lm.make_opts(validate_level=1, timing=1, round_loop=a.round_loop, key_cache=int(a.key_cache))
h = lm.lmatch_create_device(dg.offsets, dg.col, dg.w, dg.n, dg.m, opts, stream)
n = dg.n
dg = None
torch.cuda.empty_cache()
d_mate = torch.empty(max(1, n), dtype=torch.int32, device=dev)
for r in range(a.runs):
    st = lm.lmatch_run_device(h, d_mate, stream)
    print(f"run {r}: rounds={st.rounds} ms_total={st.ms_total:.3f} sweep={st.ms_sweep:.3f} "
          f"r1rest={st.ms_round1_rest:.3f} rounds_ms={st.ms_rounds:.3f} fin={st.ms_finish:.3f}", flush=True)
lm.lmatch_destroy(h)
