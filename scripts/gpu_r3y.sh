F=gpurun_out/r3y; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
for i in 1 2; do for pr in 1 2 4; do timeout 200 python bench.py --workload tdes --quick --no-configs --producers $pr 2>/dev/null | tail -1 > $F/tdes_p${pr}_$i.json; done; done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
