# Bench lines of every config + GPU tests + smoke + BB timelines (no ncu):
# the part of scripts/measure_final.sh that changes with host-side / buffer changes
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/gputest.txt 2>&1; echo gputest=$?; tail -2 gpurun_out/gputest.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; echo smoke=$?
timeout 900 python bench.py > gpurun_out/r02_bench_bb.json 2> gpurun_out/r02_bench_bb.err; echo bb=$?
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r02_bench_ref.json 2> gpurun_out/r02_bench_ref.err
for c in tiny bl vt; do timeout 900 python bench.py --config $c > gpurun_out/r02_bench_$c.json 2> gpurun_out/r02_bench_$c.err; echo $c=$?; done
timeout 1200 python bench.py --config lm > gpurun_out/r02_bench_lm.json 2> gpurun_out/r02_bench_lm.err; echo lm=$?
timeout 1200 python bench.py --config l8 > gpurun_out/r02_bench_l8.json 2> gpurun_out/r02_bench_l8.err; echo l8=$?
timeout 900 python bench.py --config lm --decode-steps 4 --steps 3 --no-cpu > gpurun_out/r02_bench_lm_decode4.json 2> gpurun_out/r02_bench_lm_decode4.err
timeout 600 python bench.py --config bbp --no-cpu > gpurun_out/r02_bench_bbp.json 2> gpurun_out/r02_bench_bbp.err
timeout 600 python bench.py --plan cut6 --no-cpu > gpurun_out/r02_bench_bb_cut6.json 2> gpurun_out/r02_bench_bb_cut6.err
timeout 300 python scripts/timeline.py bb 1 3 > gpurun_out/r02_timeline_bb_layer.txt 2>&1
timeout 300 python scripts/pipeline_timeline.py bb 4096 10 4 > gpurun_out/r02_pipeline_timeline_bb.txt 2>&1
for f in gpurun_out/r02_bench_*.json; do python -c "import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', d.get('value'), d.get('unit'), d.get('ms_per_step'), (d.get('roofline') or {}).get('frac'), (d.get('clocks') or {}).get('sm_mhz'))" 2>/dev/null; done
