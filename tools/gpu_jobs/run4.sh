cd $GRAFT_REPO_ROOT
python -m pytest tests/test_gpu_parity.py -q -k "k2_cluster or overflow or precision" > gpurun_out/t4.log 2>&1; echo rc=$? >> gpurun_out/t4.log
tail -3 gpurun_out/t4.log
python tools/k2_timing.py
SW_K2_BIG=1000000000000 python tools/k2_timing.py
python tools/k2_timing.py --m 30000 --n 20000 --reps 2
SW_K2_BIG=1000000000000 python tools/k2_timing.py --m 30000 --n 20000 --reps 2
python tools/c5_tail.py --n-db 256 --reps 3
python tools/c5_tail.py --n-db 512 --reps 3
