F=gpurun_out/r2q; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_bruteforce.py tests/test_gpu_runtime.py tests/test_gpu_parity.py -m gpu -q -x -k "not full_size" > $F/pytest.log 2>&1
bash scripts/build_variants.sh hpl "-DPAGODA_LOOKAHEAD=2 -DPAGODA_CLAIM_SMALL=2" > $F/variants.log 2>&1
VARS="0 hpl" AB=r2q ABW="tdes mm nop mb" bash scripts/gpu_ab.sh > $F/ab.txt 2>&1
tail -2 $F/pytest.log; cat $F/ab.txt
