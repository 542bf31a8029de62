python -m paper_conf_sc_abdelfattahgbtld22_b200.build > gpurun_out/ea_build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_extend_add.py -q > gpurun_out/pytest_ea.log 2>&1; echo pytest rc $?; tail -3 gpurun_out/pytest_ea.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 300 python tools/bench_extend_add.py > gpurun_out/bench_ea.json 2> gpurun_out/bench_ea.err; cat gpurun_out/bench_ea.json; tail -3 gpurun_out/bench_ea.err
timeout 300 python tools/bench_extend_add.py --parents 8192 --np-max 256 > gpurun_out/bench_ea_small.json 2>> gpurun_out/bench_ea.err; cat gpurun_out/bench_ea_small.json
timeout 600 ncu --set full --clock-control none -k regex:extend_add -c 2 -o gpurun_out/prof_ea python tools/bench_extend_add.py --reps 1 > gpurun_out/ncu_ea.log 2>&1; tail -1 gpurun_out/ncu_ea.log
