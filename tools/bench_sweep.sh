#!/bin/bash
# bench_sweep.sh "<label>|<VAR=val ...>|<bench args>" ... : short C4 bench lines for tuning experiments
# (3 timed steps, no e2e / cpu baseline), one summary line per setting into gpurun_out/sweep.txt
mkdir -p gpurun_out
for spec in "$@"; do
  IFS='|' read -r label envs args <<< "$spec"
  env $envs python bench.py $args --steps 3 --warmup 2 --e2e-steps 0 --no-cpu-baseline > gpurun_out/sweep_$label.log 2>&1
  python - "$label" <<'PY' >> gpurun_out/sweep.txt
import json, sys
lab = sys.argv[1]
try:
    d = json.loads(open(f"gpurun_out/sweep_{lab}.log").read().strip().splitlines()[-1])
    r = d["roofline"]
    print(f"{lab:24s} {d['value']:8.1f} GCUPS  frac {r['frac']:.3f}  k1_alone {r['k1_alone_gcups'] or 0:7.1f}  "
          f"k3_alone {r['k3_alone_gcups'] or 0:7.1f}  units {d['config']['units_per_step']}  clk {d['clocks']['sm_mhz']}")
except Exception as e:
    print(f"{lab:24s} FAILED {e}")
PY
done
