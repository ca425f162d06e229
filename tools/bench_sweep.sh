#!/bin/bash
# Parameter sweep on the bench workload: each line is "label ENV=..." ; prints value and the
# K1-alone roofline fraction.  Usage: tools/bench_sweep.sh "base" "w2 SW_K1_WAVES=2" ...
for spec in "$@"; do
  label=${spec%% *}; envs=${spec#* }; [ "$envs" = "$spec" ] && envs=""
  line=$(env $envs python bench.py --steps ${STEPS:-3} --warmup 2 --e2e-steps 0 --no-cpu-baseline ${BENCH_ARGS:-} 2>/dev/null | tail -1)
  python - "$label" "$line" <<'PY'
import json, sys
d = json.loads(sys.argv[2]); r = d["roofline"]
print(f'{sys.argv[1]:12s} step {d["value"]:8.1f} GCUPS  k1_alone {r["achieved"]:8.1f} (frac {r["frac"]:.3f})  units {d["config"]["units_per_step"]}  k3_alone {r["k3_alone_gcups"]:.0f}', flush=True)
PY
done
