for m in 8 12 10; do
  touch paper_conf_sc_abdelfattahgbtld22_b200/csrc/getrs_vec.cu
  IRR_NVCC_EXTRA="-DGV_MINB=$m" python -m paper_conf_sc_abdelfattahgbtld22_b200.build > gpurun_out/build_$m.log 2>&1
  for args in "--nrhs 1" "--batch 2000 --n-max 1024 --nrhs 1"; do echo "minb=$m $(timeout 300 python tools/bench_getrs.py $args 2>&1 | tail -1)"; done
done | tee gpurun_out/bench_getrs_minb.txt
