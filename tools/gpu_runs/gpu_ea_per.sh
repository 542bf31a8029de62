for v in 16384 4096 65536; do
  touch paper_conf_sc_abdelfattahgbtld22_b200/csrc/extend_add.cu
  IRR_NVCC_EXTRA="-DEA_PER_CTA=$v" python -m paper_conf_sc_abdelfattahgbtld22_b200.build > gpurun_out/build_$v.log 2>&1; tail -2 gpurun_out/build_$v.log
  for args in "" "--parents 8192 --np-max 256" "--parents 65536 --np-max 64"; do echo "per=$v $(timeout 300 python tools/bench_extend_add.py $args 2>&1 | tail -1)"; done
done | tee gpurun_out/bench_ea_per.txt
