# Round-end measurement pass (run on the GPU box from the repo root):
# bench lines for every config, the ncu launch list of the BB bench command
# and one --set full capture of a BB split run.
set -x
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_bb.json 2> gpurun_out/bench_bb.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for c in tiny bl vt lm; do python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; done
python bench.py --plan cut6 --no-cpu > gpurun_out/bench_bb_cut6.json 2> gpurun_out/bench_bb_cut6.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_bb.csv python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on \
  -k regex:"gemm_bf16|attn_tc|ramp_bert|ln_compact|layernorm_kernel|gemm_ln" -c 10 \
  -o gpurun_out/layer_full python scripts/layer_time.py 1 > gpurun_out/ncu_full.log 2>&1
