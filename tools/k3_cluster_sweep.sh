#!/bin/bash
# sweep K3 cluster sizes
cd $GRAFT_REPO_ROOT
python -m pytest tests/test_gpu_parity.py -m gpu -q -k "cluster_split" > gpurun_out/sweep_tests.log 2>&1; echo rc=$? >> gpurun_out/sweep_tests.log
run() { label=$1; shift; line=$(env "$@" python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline $BARGS 2>/dev/null | tail -1); python -c "
import json,sys; d=json.loads(sys.argv[2]); print(sys.argv[1], round(d['value'],1), d['config'].get('units_per_step'), flush=True)" "$label" "$line"; }
for c in 0 3 4 5 8; do BARGS="--config C5 --n-db 256" run "C5@256 C=$c" SW_K3_CLUSTER=$c; done
for c in 0 3 4 5; do BARGS="--config C5 --n-db 512" run "C5@512 C=$c" SW_K3_CLUSTER=$c; done
for c in 4 5 3; do BARGS="--config C4 --n-db 67188" run "C4@1/8 mixc=$c" SW_K3_MIXC=$c; done
