# Same-box A/B of a diagnostics environment switch on bench configs:
# bash scripts/ab_env.sh "E3_ATTN_STATIC=1" bb vt   (runs base, variant, base, variant)
v="$1"; shift
for rep in 1 2; do
  echo "== base"; bash scripts/quick_bench.sh "$@"
  echo "== $v"; env $v bash scripts/quick_bench.sh "$@"
done
