export MOBIUS_KT_NOSYNC=1
for i in 1 2; do
python tools/gemm_epi_ab.py 32768 6400 1600 0 2
for v in MOBIUS_EPI_NOGELU1 MOBIUS_EPI_NOAUX1 MOBIUS_EPI_NOAUX1_MOBIUS_EPI_NOGELU1; do echo $v; MOBIUS_LIB_PATH=tools/gpu/var/libmobius_$v.so python tools/gemm_epi_ab.py 32768 6400 1600 2; done
done
