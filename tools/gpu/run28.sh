export MOBIUS_KT_NOSYNC=1
python tools/gemm_epi_ab.py 32768 6400 1600 0 1 2 4
python tools/gemm_epi_ab.py 32768 1600 1600 0 1 3
python tools/gemm_epi_ab.py 32768 4800 1600 0 1
python tools/gemm_epi_ab.py 32768 6400 1600 0 1 2 4
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc2 -s 3 -c 1 -o gpurun_out/fc1_gelu python tools/gemm_one.py 32768 6400 1600 0 1 2 0 -1 -1 5 > gpurun_out/fc1ncu.log 2>&1; echo ncu rc=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc2 -s 3 -c 1 -o gpurun_out/fc1_plain python tools/gemm_one.py 32768 6400 1600 0 1 0 0 -1 -1 5 >> gpurun_out/fc1ncu.log 2>&1; echo ncu rc=$?
