F=gpurun_out/r2i; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh nolf "-DPAGODA_LOCAL_FIT=0" > $F/variants.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bruteforce.py -m gpu -q -x -k "mb or mandel or brute or ledger or mm" > $F/pytest.log 2>&1
VARS="0 nolf" AB=r2i ABW="mb tdes mm nop" bash scripts/gpu_ab.sh > $F/ab.txt 2>&1
for m in 1 2; do timeout 200 python bench.py --workload mm --quick --no-configs --mtbs $m --arena-kb 64 2>/dev/null | tail -1 > $F/mm_m$m.json; python -c "import json;d=json.loads(open('$F/mm_m$m.json').read());print('mm m$m', round(d['value']/1e6,2))" >> $F/ab.txt; done
tail -3 $F/pytest.log; cat $F/ab.txt
