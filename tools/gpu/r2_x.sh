# round 2, session X: shorter dependent chains (apply V2 grow reservations in one atomic round, M12 stamps/records
# preloaded, F0 pending count + F1 psi0 marks folded into the filter / commit passes): full GPU suite, A/B vs base
set -x
mkdir -p gpurun_out
AB=$PWD/paper_conf_dac_leejlczcshh25_b200/ab
timeout 1700 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/x_pytest.txt 2>&1
tail -3 gpurun_out/x_pytest.txt
for rep in 1 2; do
for v in main base; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 400 python bench.py --steps 40 --no-cpu-baseline --no-repartition > gpurun_out/x_bench_c2_${v}_$rep.json 2> gpurun_out/x_bench_c2_${v}_$rep.err
done
done
for v in main base; do
  if [ $v = main ]; then L=""; else L="IGK_LIB=$AB/libigk_$v.so"; fi
  env $L timeout 500 python bench.py --config C4 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/x_bench_c4_$v.json 2> gpurun_out/x_bench_c4_$v.err
  env $L timeout 500 python bench.py --config C5 --steps 10 --no-cpu-baseline --no-repartition > gpurun_out/x_bench_c5_$v.json 2> gpurun_out/x_bench_c5_$v.err
done
IGK_FLUSH=1 IGK_DEBUG_ARRIVALS=1 timeout 300 python tools/phase_profile.py 12 C2 > gpurun_out/x_phase_c2.txt 2>&1
for f in gpurun_out/x_bench_*.json; do echo $f; python -c "import json,sys; d=json.loads(open('$f').read().strip().split(chr(10))[-1]); print(d['ms_per_step'], d['iteration']['ms_p50'], d['e2e']['ms_per_step'], d['roofline_s9']['launch_ms'])"; done
