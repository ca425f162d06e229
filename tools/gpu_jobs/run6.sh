cd $GRAFT_REPO_ROOT
python -m pytest tests -m gpu -x -q > gpurun_out/t6.log 2>&1; echo rc=$? >> gpurun_out/t6.log
tail -3 gpurun_out/t6.log
python tools/k2_timing.py
python tools/k2_timing.py --m 30000 --n 20000 --reps 2
python tools/k2_timing.py --m 10000 --n 20000 --reps 2
SW_K2_BIG=1000000000000 python tools/k2_timing.py --m 10000 --n 20000 --reps 2
python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline --config C5 --n-db 256 | tail -1 | cut -c 1-200
python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu-baseline | tail -1 | cut -c 1-200
