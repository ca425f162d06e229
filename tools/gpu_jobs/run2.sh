cd $GRAFT_REPO_ROOT
python -m pytest tests/test_gpu_parity.py -q -k "k2_cluster or overflow or precision or cluster_split" > gpurun_out/t2.log 2>&1; echo rc=$? >> gpurun_out/t2.log
tail -3 gpurun_out/t2.log
python tools/k2_timing.py
SW_K2_BIG=1000000000000 python tools/k2_timing.py
run() { label=$1; shift; line=$(env "$@" python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline $BARGS 2>/dev/null | tail -1); python -c "
import json,sys; d=json.loads(sys.argv[2]); print(sys.argv[1], round(d['value'],1), d['config'].get('units_per_step'), d['config'].get('overflow_pairs'), flush=True)" "$label" "$line"; }
BARGS="--config C5 --n-db 256" run "C5@256 new" X=1
BARGS="--config C5 --n-db 256" run "C5@256 k2single" SW_K2_BIG=1000000000000
BARGS="--config C5 --n-db 512" run "C5@512 new" X=1
BARGS="--config C5" run "C5 new" X=1
BARGS="--config C4 --n-db 67188" run "C4@1/8 new" X=1
