# cold bodies behind calls in the 4-MTB/SM kernel
F=gpurun_out/r4g; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_parity.py -q -x -k "four or mm or mandelbrot" > $F/pytest.log 2>&1; tail -2 $F/pytest.log
PAGODA_TEST_FLAGS=0x40 timeout 600 python -m pytest tests/test_gpu_workloads.py -q -x -k "c5 or mix" > $F/pytest_w.log 2>&1; tail -2 $F/pytest_w.log
for i in 1 2; do for w in mm mm_tc mm_noshm tdes mb; do timeout 200 python bench.py --workload $w --quick --no-configs 2>/dev/null | tail -1 > $F/${w}_0_$i.json; done; done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
