# round 2, session H: pre-load change A/B, sanitizers re-run, apply/refine C4 ncu with source
set -x
timeout 400 python bench.py --steps 30 --no-cpu-baseline --no-repartition > gpurun_out/h_bench_c2.json 2> gpurun_out/h_bench_c2.err
timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/h_bench_c4.json 2> gpurun_out/h_bench_c4.err
for t in racecheck initcheck; do
  timeout 900 compute-sanitizer --tool $t python tools/sanitize_c1.py > gpurun_out/h_san_$t.txt 2>&1
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_apply|k_refine" -s 5 -c 2 -o gpurun_out/h_split_c4 python tools/profile_step.py C4 4 > gpurun_out/h_ncu.log 2>&1
timeout 1700 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/h_pytest.txt 2>&1
for f in gpurun_out/h_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['value'])"; done
tail -2 gpurun_out/h_san_*.txt gpurun_out/h_pytest.txt
