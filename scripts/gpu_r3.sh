python -c "import __graft_entry__ as g; g.build()" > /dev/null
timeout 300 python scripts/probe_runtime.py > gpurun_out/probe_runtime.json 2>&1
for w in mm tdes; do timeout 300 python bench.py --workload $w --prespawn --quick --no-cpu --no-naive --steps 5 > gpurun_out/pre_$w.json 2>&1; done
export PAGODA_LIB=$PWD/build/variants/libpagoda_v1.so
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "tdes and not naive" 2>&1 | tail -1 > gpurun_out/var_t1.txt
for i in 1 2 3; do timeout 300 python bench.py --workload tdes --quick --no-cpu --no-naive 2>/dev/null | tail -1 > gpurun_out/var_b1_$i.json; done
unset PAGODA_LIB
for i in 1 2 3; do timeout 300 python bench.py --workload tdes --quick --no-cpu --no-naive 2>/dev/null | tail -1 > gpurun_out/var_b0_$i.json; done
timeout 300 python -m pytest tests/test_gpu_runtime.py -q -x -k pingpong 2>&1 | tail -1 > gpurun_out/pp_test.txt
timeout 900 python scripts/sweeps.py > gpurun_out/sweeps.jsonl 2> gpurun_out/sweeps.err
