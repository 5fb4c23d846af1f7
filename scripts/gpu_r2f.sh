F=gpurun_out/r2f; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh old "-DPAGODA_FAST_LOAD=0 -DPAGODA_FAST_PUB=0" > $F/variants.log 2>&1
timeout 600 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py -m gpu -q -x > $F/pytest.log 2>&1
VARS="0 old" AB=r2f ABW="tdes mm nop mb mix" bash scripts/gpu_ab.sh > $F/ab.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master_kernel -c 1 -o $F/ncu_tdes python bench.py --quick --no-configs --prespawn --steps 1 --warmup 0 > $F/ncu_run.log 2>&1
tail -2 $F/pytest.log; cat $F/ab.txt
