# round 2 (session 2) evidence run -> gpurun_out/final2 (copied to profiles/r02/final2)
export PATH=/usr/local/cuda/bin:$PATH
O=gpurun_out/final2; mkdir -p $O
nvidia-smi --query-gpu=name,driver_version,clocks.max.sm --format=csv > $O/smi.txt; lscpu | grep 'Model name' >> $O/smi.txt; nproc >> $O/smi.txt; free -g >> $O/smi.txt
( time timeout 1800 python -m pytest tests -q -m gpu -s -p no:randomly ) > $O/pytest_gpu.log 2>&1; echo pytest rc $?; tail -4 $O/pytest_gpu.log; grep "\[parity" $O/pytest_gpu.log | cut -c1-200
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke rc $?; tail -1 $O/smoke.log
timeout 900 python bench.py > $O/bench_default_C5.json 2> $O/bench_default_C5.err; echo bench rc $?; tail -c 2500 $O/bench_default_C5.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference_C5.json 2>&1; echo ref rc $?; tail -c 400 $O/bench_reference_C5.json
for c in C1big C2 C3; do timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; echo "$c rc $?"; done
timeout 600 python bench.py --config C4 --steps 3 > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc $?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C5.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu-launch rc $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:xgemm_ws -s 3 -c 1 -o $O/prof_xgemm_C5 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > $O/ncu_xgemm.log 2>&1; echo ncu-full rc $?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:outer_swap_trsm -s 3 -c 1 -o $O/prof_outer_C5 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > $O/ncu_outer.log 2>&1; echo ncu-full2 rc $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:lu_small_kernel -c 4 -o $O/prof_small_C1big python tools/prof_one.py --config C1big --reps 1 > $O/ncu_small.log 2>&1; echo ncu-small rc $?
for w in tierS grid2 partial; do
  for t in memcheck racecheck synccheck; do
    timeout 600 compute-sanitizer --tool $t --print-limit 10 python tools/sanitize_run.py $w > $O/san_${w}_${t}.log 2>&1
    echo "$w $t rc=$? $(grep -h 'ERROR SUMMARY\|RACECHECK SUMMARY' $O/san_${w}_${t}.log | tr '\n' ' ')"
  done
done
timeout 900 python tools/bench_next.py --reps 3 > $O/bench_next.jsonl 2> $O/bench_next.err; echo next rc $?
