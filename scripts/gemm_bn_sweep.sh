C="8192,3072,768,bias_gelu 8192,3072,768,bias 8192,768,3072,bias_resid 8192,768,768,bias_resid 8192,2304,768,bias"
for bn in 0 256 192 128; do echo "BN=$bn"; E3_GEMM_BN=$bn python scripts/gemm_sweep.py $C; done
