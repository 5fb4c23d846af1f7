F=gpurun_out/r2n; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
bash scripts/build_variants.sh crel "-DPAGODA_CELL_RELAXED=1" e24 "-DPAGODA_CLAIM_SMALL=2" > $F/variants.log 2>&1
timeout 900 python -m pytest tests/test_gpu_bruteforce.py -m gpu -q -x > $F/pytest.log 2>&1
VARS="0 crel" AB=r2n ABW="tdes mm nop" bash scripts/gpu_ab.sh > $F/ab.txt 2>&1
for ew in 16 24; do timeout 200 python bench.py --quick --no-configs --exec-warps $ew 2>/dev/null | tail -1 > $F/tdes_ew$ew.json; python -c "import json;d=json.loads(open('$F/tdes_ew$ew.json').read());print('tdes ew$ew', round(d['value']/1e6,2))" >> $F/ab.txt; done
tail -3 $F/pytest.log; cat $F/ab.txt
