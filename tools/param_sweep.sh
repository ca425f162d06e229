set -u
mkdir -p gpurun_out/sweep
timeout 400 python bench.py --config C5 > gpurun_out/sweep/c5.log 2>&1
for s in 3 4 6 8; do timeout 200 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 --streams $s > gpurun_out/sweep/c4_s$s.log 2>&1; done
for lt in 2048 4096 6144; do timeout 200 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 --long-threshold $lt > gpurun_out/sweep/c4_lt$lt.log 2>&1; done
for uc in 25000000000 100000000000 200000000000; do timeout 200 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 --unit-cells $uc > gpurun_out/sweep/c4_uc$uc.log 2>&1; done
for f in gpurun_out/sweep/*.log; do echo $f $(grep '^{' $f | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print(round(d['value'],1), d['config'].get('units_per_step'), d['config'].get('streams_per_gpu'))" 2>&1); done
