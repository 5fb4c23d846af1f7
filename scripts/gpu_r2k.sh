F=gpurun_out/r2k; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_bruteforce.py tests/test_gpu_parity.py tests/test_gpu_runtime.py -m gpu -q -x -k "brute or two_scheduling or ledger or nop_many or mark or barrier or single_mtb or spread or four" > $F/pytest.log 2>&1
for g in 1 2; do for i in 1 2; do
  timeout 200 python bench.py --quick --no-configs --groups $g 2>/dev/null | tail -1 > $F/tdes_g${g}_$i.json
  timeout 200 python bench.py --quick --no-configs --workload nop --groups $g 2>/dev/null | tail -1 > $F/nop_g${g}_$i.json
  timeout 200 python bench.py --quick --no-configs --workload mm --groups $g --mtbs 2 --arena-kb 64 2>/dev/null | tail -1 > $F/mm2_g${g}_$i.json
  timeout 200 python bench.py --quick --no-configs --workload mix --groups $g 2>/dev/null | tail -1 > $F/mix_g${g}_$i.json
done; done
for f in $F/*.json; do python -c "import json;d=json.loads(open('$f').read());print('$f', round(d['value']/1e6,2), round(d['roofline']['frac'] or 0,3))" 2>/dev/null || echo "$f failed"; done > $F/summary.txt
tail -3 $F/pytest.log; cat $F/summary.txt
