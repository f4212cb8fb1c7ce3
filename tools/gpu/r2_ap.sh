# round 2, session AP: validation of the final HEAD (65c5a1f): full GPU suite, smoke, default bench, launch list
set -x
mkdir -p gpurun_out
timeout 1700 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/ap_pytest.txt 2>&1
tail -3 gpurun_out/ap_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/ap_smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/ap_bench_c2.json 2> gpurun_out/ap_bench_c2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/ap_launches_c2.csv python bench.py --steps 3 --warmup 3 --profile > /dev/null 2>&1
cat gpurun_out/ap_smoke.txt; tail -c 600 gpurun_out/ap_bench_c2.json
