# bench lines for every config (no profilers), into gpurun_out/bench_<cfg>.json
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_bb.json 2> gpurun_out/bench_bb.err
python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for c in tiny bl vt lm; do python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; done
python bench.py --plan cut6 --no-cpu > gpurun_out/bench_bb_cut6.json 2> gpurun_out/bench_bb_cut6.err
