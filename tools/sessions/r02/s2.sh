M=gpurun_out/s2; mkdir -p $M
timeout 600 python -m pytest tests/test_gpu_multirank.py -x -q -k "query or watchdog or collectives" > $M/pytest_comm.log 2>&1; echo "comm rc=$?"; tail -5 $M/pytest_comm.log
timeout 300 python bench.py --gpus 2 --steps 2 > $M/gpus2.log 2>&1; echo "gpus2 rc=$?"; tail -2 $M/gpus2.log
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"; tail -c 600 $M/bench_default.log
