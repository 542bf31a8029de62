python -m paper_conf_sc_abdelfattahgbtld22_b200.build > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_extend_add.py -q > gpurun_out/pytest_ea.log 2>&1; echo pytest rc $?; tail -15 gpurun_out/pytest_ea.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
for args in "" "--parents 8192 --np-max 256" "--parents 65536 --np-max 64" "--parents 65536 --np-max 85"; do echo "$(timeout 300 python tools/bench_extend_add.py $args 2>&1 | tail -1)"; done | tee gpurun_out/bench_ea_small_kernel.txt
