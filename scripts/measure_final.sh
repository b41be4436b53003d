# End-of-round measurement pass (on the GPU box, from the repo root): GPU
# tests, smoke, bench lines for every config, device timelines, kernel
# micro-benchmarks, the ncu launch list of the BB bench command, one --set
# full capture of a BB split run, and compute-sanitizer on the tiny pipelines.
# Outputs under gpurun_out/ (copied into profiles/ as r02_* by the builder).
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gputest.txt 2>&1; echo gputest=$?; tail -2 gpurun_out/gputest.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; echo smoke=$?
timeout 900 python bench.py > gpurun_out/r02_bench_bb.json 2> gpurun_out/r02_bench_bb.err; echo bb=$?
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r02_bench_ref.json 2> gpurun_out/r02_bench_ref.err
for c in tiny bl vt; do timeout 900 python bench.py --config $c > gpurun_out/r02_bench_$c.json 2> gpurun_out/r02_bench_$c.err; echo $c=$?; done
timeout 1200 python bench.py --config lm > gpurun_out/r02_bench_lm.json 2> gpurun_out/r02_bench_lm.err; echo lm=$?
timeout 900 python bench.py --config lm --decode-steps 4 --steps 3 --no-cpu > gpurun_out/r02_bench_lm_decode4.json 2> gpurun_out/r02_bench_lm_decode4.err
timeout 600 python bench.py --config bbp --no-cpu > gpurun_out/r02_bench_bbp.json 2> gpurun_out/r02_bench_bbp.err
timeout 600 python bench.py --plan cut6 --no-cpu > gpurun_out/r02_bench_bb_cut6.json 2> gpurun_out/r02_bench_bb_cut6.err
timeout 300 python scripts/timeline.py bb 1 3 > gpurun_out/r02_timeline_bb_layer.txt 2>&1
timeout 300 python scripts/pipeline_timeline.py bb 4096 10 4 > gpurun_out/r02_pipeline_timeline_bb.txt 2>&1
timeout 300 python scripts/llama_timeline.py 4 > gpurun_out/r02_timeline_llama_layers.txt 2>&1
timeout 300 python scripts/dec_bench.py > gpurun_out/r02_dec_bench.txt 2>&1
(timeout 120 python scripts/attn_bench.py; timeout 120 python scripts/attn_bench.py 256 197 768 12) > gpurun_out/r02_attn_bench.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_bb.csv python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e --inputs-per-gpu 2048 > gpurun_out/ncu_bench.log 2>&1; echo ncu1=$?
timeout 1200 ncu --set full --clock-control none --import-source on \
  -k regex:"gemm_bf16|attn_tc|ramp_bert|ln_compact|layernorm_kernel|gemm_ln" -c 10 \
  -o gpurun_out/layer_full python scripts/layer_time.py 1 > gpurun_out/ncu_full.log 2>&1; echo ncu2=$?
for t in memcheck synccheck; do
  echo "# compute-sanitizer --tool $t --print-limit 40 python scripts/sanitize_run.py   (B200, end of round 2; tiny BERT / tiny ViT / tiny LLaMA bf16 + FP32, 2-rank LOOPBACK stage pipeline)" > gpurun_out/san_$t.txt
  timeout 1500 compute-sanitizer --tool $t --print-limit 40 python scripts/sanitize_run.py >> gpurun_out/san_$t.txt 2>&1; echo $t=$?
done
for f in gpurun_out/r02_bench_*.json; do python -c "import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d.get('value'), d.get('unit'), d.get('ms_per_step'), (d.get('roofline') or {}).get('frac'), (d.get('clocks') or {}).get('sm_mhz'))" 2>/dev/null; done
