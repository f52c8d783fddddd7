export MOBIUS_KT_NOSYNC=1 GEMM_T=32768
python tools/gemm_prof.py && \
timeout 900 ncu --set full --kernel-name regex:gemm_tc2 -c 12 -o gpurun_out/r3_gemm_full python tools/gemm_prof.py > gpurun_out/r3_gemm_ncu.log 2>&1; echo rc=$?
