export PAGODA_LIB=$PWD/build/variants/libpagoda_vimad.so
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_workloads.py -q -x -k "tdes or mpe" 2>&1 | tail -1
for r in 1 2 3; do for v in 0 imad; do
  if [ $v = 0 ]; then unset PAGODA_LIB; else export PAGODA_LIB=$PWD/build/variants/libpagoda_v$v.so; fi
  timeout 300 python bench.py --workload tdes --quick --no-cpu --no-naive --steps 10 2>/dev/null | tail -1 > gpurun_out/ab10_${v}_$r.json
  echo "$v $r $(python -c "import json;d=json.load(open('gpurun_out/ab10_${v}_$r.json'));print(round(d['value']/1e6,3), round(d['roofline']['frac'],3))")"
done; done
export PAGODA_LIB=$PWD/build/variants/libpagoda_vimad.so
timeout 900 ncu --set full --clock-control none -k regex:master -s 3 -c 1 -o gpurun_out/tdes_imad \
  python bench.py --workload tdes --prespawn --steps 1 --warmup 3 --no-naive --no-cpu --quick > /dev/null 2>&1
python scripts/ncu_summary.py gpurun_out/tdes_imad.ncu-rep > gpurun_out/ncu_tdes_imad.txt 2>&1; rm -f gpurun_out/tdes_imad.ncu-rep; head -16 gpurun_out/ncu_tdes_imad.txt
