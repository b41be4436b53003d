set -x
for m in 0 1 2 4 8 16 32 64 128 192; do echo "SKIP=$m"; E3_SKIP=$m python scripts/layer_time.py 1 2>&1 | tail -1; done > gpurun_out/knockout.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"gemm_bf16_tc_kernel|ramp_bert|ln_compact|layernorm_kernel|attn_tc" -c 8 -o gpurun_out/layer_full python scripts/layer_time.py 1 > gpurun_out/ncu_layer.log 2>&1
