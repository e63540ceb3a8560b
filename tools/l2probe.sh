python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for n in 4000000 8000000 16000000 32000000 64000000 128000000; do
python bench.py --n $n --steps 20 --warmup 5 --no-e2e --no-cpu-baseline 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.load(sys.stdin); s=d['stages_ms_per_step']; n=$n
print(n, 'step %.3f'%d['ms_per_step'], ' '.join('%s=%.3f'%(k, v*1e9/n) for k,v in s.items() if k.startswith('sort') or k=='prepass'), 'passes', d['config']['sort_passes'])"
done
python tools/distinct_probe.py C5 > gpurun_out/distinct_c5.txt 2>&1
