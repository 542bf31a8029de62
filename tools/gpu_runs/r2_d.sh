export PATH=/usr/local/cuda/bin:$PATH
for s in "8192x700" "5000x3000" "3000x5000" "4096x4096"; do
  timeout 300 compute-sanitizer --tool memcheck --print-limit 5 python tools/repro_large.py $s > gpurun_out/san_$s.log 2>&1; echo "$s rc $?"; grep -E "Invalid|ok|ERROR|Error" gpurun_out/san_$s.log | head -8
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C3_outer.csv python bench.py --config C3 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --tune nb_outer=128 > /dev/null 2>&1; echo ncu1 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:outer_swap_trsm -s 20 -c 2 -o gpurun_out/prof_outer_trsm_C3 python bench.py --config C3 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --tune nb_outer=128 > gpurun_out/ncu_outer.log 2>&1; echo ncu2 $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:xgemm_sched -s 20 -c 2 -o gpurun_out/prof_xgemm_C3 python bench.py --config C3 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --tune nb_outer=128 > gpurun_out/ncu_xgemm.log 2>&1; echo ncu3 $?
