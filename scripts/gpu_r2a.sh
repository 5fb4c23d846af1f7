set -x
F=gpurun_out/r2a; mkdir -p $F
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $F/smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $F/smoke.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $F/smoke_launches.csv python -c "import __graft_entry__ as g; g.smoke()" > $F/smoke_ncu.log 2>&1
timeout 900 python -m pytest tests/test_gpu_bruteforce.py tests/test_gpu_runtime.py tests/test_cpp_api.py -m gpu -q -x -s > $F/pytest_new.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $F/pytest_gpu.log 2>&1
tail -5 $F/pytest_new.log $F/pytest_gpu.log
