#!/bin/bash
# Run bench + a quick parity check for every variant in build/variants (builder tooling; GPU box).
cd "$(dirname "$0")/.."
for f in build/variants/*.so; do
  LMATCH_LIB=$PWD/$f python - <<'PY'
import os, sys, numpy as np
sys.path.insert(0, os.getcwd())
import graphgen, oracle, paper_conf_sc_mandulakgfhs24_b200 as lm
ok = True
for g in (graphgen.rmat(16, 16, seed=3), graphgen.mesh(200, keep=0.6, seed=2), graphgen.er(20000, 3.0, seed=1)):
    with lm.Matcher(g) as M:
        mate, st = M.run()
    ok &= bool(np.array_equal(mate, oracle.greedy(g).mate))
print(os.path.basename(os.environ["LMATCH_LIB"]), "parity", ok, flush=True)
PY
  for wl in "rmat --scale 26" "road --scale 26" "gradient --scale 18"; do
    LMATCH_LIB=$PWD/$f python bench.py --workload $wl --no-e2e --no-cpu --steps 10 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read())
print('   ', d['config']['workload'][:12], 'GTEPS %.2f' % d['value'], 'step %.3f ms' % d['ms_per_step'], 'sweep %.3f ms frac %.3f' % (d['roofline']['launch_ms'], d['roofline']['frac']), flush=True)"
  done
done
