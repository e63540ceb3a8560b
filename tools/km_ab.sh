# k-means option: compile-time variants on C5 (k = 3)
for defs in "$@"; do
  SR_EXTRA_NVCC="$defs" python -c "import paper_conf_micro_chungnkk25_b200 as s; s.build(force=True)" || continue
  echo -n "[$defs] "; python bench.py --split 3 --steps 2 --warmup 1 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "import json,sys; d=json.load(sys.stdin); print(d['ms_per_step'])"
done
python -c "import paper_conf_micro_chungnkk25_b200 as s; s.build(force=True)"
