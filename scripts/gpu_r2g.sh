F=gpurun_out/r2g; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh nob "-DPAGODA_BATCH_PLACE=0" fl "-DPAGODA_FAST_LOAD=1" > $F/variants.log 2>&1
timeout 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py tests/test_cpp_api.py -m gpu -q -x > $F/pytest.log 2>&1
VARS="0 nob fl" AB=r2g ABW="tdes mm nop mb mix" bash scripts/gpu_ab.sh > $F/ab.txt 2>&1
tail -3 $F/pytest.log; cat $F/ab.txt
