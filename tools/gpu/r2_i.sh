set -x
timeout 400 python bench.py --steps 30 --no-cpu-baseline --no-repartition > gpurun_out/i_bench_c2.json 2> gpurun_out/i_bench_c2.err
timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/i_bench_c4.json 2> gpurun_out/i_bench_c4.err
timeout 300 python bench.py --config C3 --k 64 --frac 0.1 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/i_bench_c3.json 2> /dev/null
timeout 400 python bench.py --config C5 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/i_bench_c5.json 2> /dev/null
timeout 400 python tools/phase_profile.py 8 C4 > gpurun_out/i_phase_c4.txt 2>&1
timeout 900 compute-sanitizer --tool initcheck python tools/sanitize_c1.py > gpurun_out/i_san_initcheck.txt 2>&1
timeout 1200 python -m pytest tests/test_gpu_paths.py tests/test_gpu_parity.py tests/test_shard.py -q -x -p no:cacheprovider -k "not 1000" > gpurun_out/i_pytest.txt 2>&1
for f in gpurun_out/i_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['value'])"; done
tail -n 3 gpurun_out/i_pytest.txt gpurun_out/i_san_initcheck.txt; cat gpurun_out/i_phase_c4.txt
