# compute-sanitizer memcheck / synccheck over scripts/sanitize_run.py and
# racecheck per config, aggregated (gpurun_out/san_*.txt)
mkdir -p gpurun_out
for t in memcheck synccheck; do
  echo "# compute-sanitizer --tool $t --print-limit 40 python scripts/sanitize_run.py   (B200, r02 end of round; tiny BERT / tiny ViT / tiny LLaMA bf16 + FP32, 2-rank LOOPBACK stage pipeline)" > gpurun_out/san_$t.txt
  timeout 1500 compute-sanitizer --tool $t --print-limit 40 python scripts/sanitize_run.py >> gpurun_out/san_$t.txt 2>&1; echo $t=$?
done
echo "# compute-sanitizer --tool racecheck --racecheck-report all, aggregated by scripts/racecheck_summary.py (B200, r02 end of round)" > gpurun_out/san_racecheck.txt
for c in tiny tiny-vit llama fp32 loopback; do
  echo "== $c" >> gpurun_out/san_racecheck.txt
  timeout 1500 compute-sanitizer --tool racecheck --racecheck-report all python scripts/sanitize_run.py $c 2>&1 | python scripts/racecheck_summary.py >> gpurun_out/san_racecheck.txt; echo race_$c=$?
done
