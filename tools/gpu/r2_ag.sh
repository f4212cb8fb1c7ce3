# round 2, session AG: final measurements of this round's build -- driver-style bench lines (C2 default,
# reference arm, C1/C3/C4/C5), ncu launch list + full capture of k_step at C2, sanitizers, smoke
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/ag_env.txt; nproc >> gpurun_out/ag_env.txt
timeout 600 python bench.py > gpurun_out/ag_bench_c2.json 2> gpurun_out/ag_bench_c2.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/ag_bench_ref.json 2> gpurun_out/ag_bench_ref.err
timeout 900 python bench.py --config C4 --steps 20 --no-cpu-baseline > gpurun_out/ag_bench_c4.json 2> gpurun_out/ag_bench_c4.err
timeout 600 python bench.py --config C5 --steps 20 --no-cpu-baseline --no-repartition > gpurun_out/ag_bench_c5.json 2> gpurun_out/ag_bench_c5.err
timeout 600 python bench.py --config C3 --k 64 --frac 0.1 --steps 20 --no-cpu-baseline --no-repartition > gpurun_out/ag_bench_c3.json 2> gpurun_out/ag_bench_c3.err
timeout 600 python bench.py --config C1 --steps 20 --no-cpu-baseline --no-repartition > gpurun_out/ag_bench_c1.json 2> gpurun_out/ag_bench_c1.err
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/ag_smoke.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/ag_launches_c2.csv python bench.py --steps 3 --warmup 3 --profile > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_step" -s 5 -c 1 -o gpurun_out/ag_step_c2 python tools/profile_step.py C2 6 > gpurun_out/ag_ncu_step.log 2>&1
for t in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $t python tools/sanitize_c1.py > gpurun_out/ag_san_$t.txt 2>&1
done
tail -2 gpurun_out/ag_san_*.txt; cat gpurun_out/ag_smoke.txt
for f in gpurun_out/ag_bench_*.json; do echo $f; tail -c 400 $f; echo; done
