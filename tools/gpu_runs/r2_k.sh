# sanitizers over every tier + the every-front C5 parity check (long)
bash tools/gpu_runs/r2_sanitize.sh 2>&1 | tee gpurun_out/sanitizer/summary.txt
IRR_PARITY_C5_ALL=1 timeout 3000 python -m pytest tests/test_gpu_fullconfig.py -q -s -p no:randomly -k c5 > gpurun_out/parity_c5_all.log 2>&1; echo c5all rc $?; grep "parity C5" gpurun_out/parity_c5_all.log; tail -2 gpurun_out/parity_c5_all.log
