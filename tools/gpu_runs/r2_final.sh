# round 2 final measurements (profiles/r02/final)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/final
nvidia-smi --query-gpu=name,driver_version,clocks.max.sm --format=csv > gpurun_out/final/smi.txt; lscpu | grep 'Model name' >> gpurun_out/final/smi.txt; nproc >> gpurun_out/final/smi.txt; free -g >> gpurun_out/final/smi.txt
( time timeout 1500 python -m pytest tests -q -m gpu -s -p no:randomly ) > gpurun_out/final/pytest_gpu.log 2>&1; echo pytest rc $?; tail -4 gpurun_out/final/pytest_gpu.log; grep "\[parity" gpurun_out/final/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final/smoke.log 2>&1; tail -1 gpurun_out/final/smoke.log
timeout 900 python bench.py > gpurun_out/final/bench_default_C5.json 2> gpurun_out/final/bench_default_C5.err; echo bench rc $?; tail -c 1500 gpurun_out/final/bench_default_C5.json
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final/bench_reference_C5.json 2>&1; echo ref rc $?; tail -c 600 gpurun_out/final/bench_reference_C5.json
for c in C1big C2 C3; do timeout 600 python bench.py --config $c > gpurun_out/final/bench_$c.json 2> gpurun_out/final/bench_$c.err; echo "$c rc $?"; done
timeout 600 python bench.py --config C4 --steps 3 > gpurun_out/final/bench_C4.json 2> gpurun_out/final/bench_C4.err; echo "C4 rc $?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/final/launches_C5.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu-launch rc $?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:xgemm_sched -s 3 -c 1 -o gpurun_out/final/prof_xgemm_C5 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/final/ncu_xgemm.log 2>&1; echo ncu-full rc $?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:outer_swap_trsm -s 3 -c 1 -o gpurun_out/final/prof_outer_C5 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/final/ncu_outer.log 2>&1; echo ncu-full2 rc $?
timeout 900 python tools/bench_next.py --reps 3 > gpurun_out/final/bench_next.jsonl 2> gpurun_out/final/bench_next.err; echo next rc $?
