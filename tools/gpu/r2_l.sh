set -x
timeout 600 python bench.py --config C4 --shard --steps 8 --no-cpu-baseline > gpurun_out/l_bench_c4_shard1.json 2> gpurun_out/l_bench_c4_shard1.err
timeout 600 python bench.py --config C4 --shard --p2p --steps 8 --no-cpu-baseline > gpurun_out/l_bench_c4_shard1_p2p.json 2> gpurun_out/l_bench_c4_shard1_p2p.err
timeout 600 python bench.py --config C2 --shard --steps 20 --no-cpu-baseline > gpurun_out/l_bench_c2_shard1.json 2> gpurun_out/l_bench_c2_shard1.err
timeout 600 python bench.py --config C2 --shard --p2p --steps 20 --no-cpu-baseline > gpurun_out/l_bench_c2_shard1_p2p.json 2> gpurun_out/l_bench_c2_shard1_p2p.err
for f in gpurun_out/l_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['value'], d['iteration']['rounds'], d['e2e']['ms_per_step'])"; done
tail -n 3 gpurun_out/l_bench_c4_shard1_p2p.err
