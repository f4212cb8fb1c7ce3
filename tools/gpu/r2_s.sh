# round 2, session S: k_recount3 (no length masks, 32-bit counters, tile prefetch) A/B vs 4 blocks/SM build;
# k_refine at 2 CTAs/SM (64 regs) A/B at C4/C3/C5; C2 per-CTA barrier arrivals with flushed L2
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
timeout 900 python -m pytest tests/test_gpu_store.py tests/test_gpu_paths.py -q -x -p no:cacheprovider > gpurun_out/s_pytest.txt 2>&1
for c in C2 C4 C5; do
  timeout 300 python tools/recount_ab.py $c 9 v3,gather > gpurun_out/s_rc_$c.txt 2>&1
  IGK_LIB=$AB/libigk_m4.so timeout 300 python tools/recount_ab.py $c 9 v3 > gpurun_out/s_rc_${c}_m4.txt 2>&1
done
timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/s_bench_c4.json 2> gpurun_out/s_bench_c4.err
IGK_LIB=$AB/libigk_rb2.so IGK_REFINE_BPS=2 timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/s_bench_c4_rb2.json 2> gpurun_out/s_bench_c4_rb2.err
timeout 500 python bench.py --config C5 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/s_bench_c5.json 2> gpurun_out/s_bench_c5.err
IGK_LIB=$AB/libigk_rb2.so IGK_REFINE_BPS=2 timeout 500 python bench.py --config C5 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/s_bench_c5_rb2.json 2> gpurun_out/s_bench_c5_rb2.err
IGK_FLUSH=1 IGK_DEBUG_ARRIVALS=1 timeout 300 python tools/phase_profile.py 30 C2 > gpurun_out/s_phase_c2.txt 2>&1
cat gpurun_out/s_rc_*.txt; tail -3 gpurun_out/s_pytest.txt
for f in gpurun_out/s_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['value'], d['roofline_s9']['launch_ms'])"; done
