# round 2, session P: full GPU suite after NEXT-2, smoke, default bench (with the GPU FGP comparator), C2 endurance 3000
set -x
timeout 1700 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/p_pytest.txt 2>&1
timeout 300 python -c "import __graft_entry__ as e; e.smoke(); print('smoke ok')" > gpurun_out/p_smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/p_bench_c2.json 2> gpurun_out/p_bench_c2.err
timeout 900 python tools/long_run.py --config C2 --iters 3000 --every 250 > gpurun_out/p_long_run_c2_3000.jsonl 2> gpurun_out/p_long_run.err
tail -n 2 gpurun_out/p_pytest.txt gpurun_out/p_smoke.txt gpurun_out/p_long_run_c2_3000.jsonl
python -c "import json; d=json.loads(open('gpurun_out/p_bench_c2.json').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['value'], d.get('full_repartition'))"
