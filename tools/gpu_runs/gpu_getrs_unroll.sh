for u in 8 16 32; do
  touch paper_conf_sc_abdelfattahgbtld22_b200/csrc/getrs_vec.cu
  IRR_NVCC_EXTRA="-DGV_UNROLL=$u" python -m paper_conf_sc_abdelfattahgbtld22_b200.build > gpurun_out/build_$u.log 2>&1
  for args in "--nrhs 1" "--batch 2000 --n-max 1024 --nrhs 1"; do echo "unroll=$u $(timeout 300 python tools/bench_getrs.py $args 2>&1 | tail -1)"; done; tail -3 gpurun_out/build_$u.log
done | tee gpurun_out/bench_getrs_unroll.txt
