python -m paper_conf_sc_abdelfattahgbtld22_b200.build > gpurun_out/build.log 2>&1; tail -2 gpurun_out/build.log
timeout 600 python -m pytest tests/test_gpu_getrs.py -q > gpurun_out/pytest_getrs.log 2>&1; echo pytest rc $?; tail -15 gpurun_out/pytest_getrs.log
for args in "--nrhs 1" "--nrhs 2" "--nrhs 4" "--nrhs 8" "--nrhs 4 --tune getrs_vec=0" "--nrhs 8 --tune getrs_vec=0" "--batch 2000 --n-max 1024 --nrhs 8" "--batch 2000 --n-max 1024 --nrhs 8 --tune getrs_vec=0"; do echo "$(timeout 300 python tools/bench_getrs.py $args 2>&1 | tail -1)"; done | tee gpurun_out/bench_getrs_r.txt
