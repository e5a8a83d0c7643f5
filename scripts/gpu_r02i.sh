#!/bin/bash
export PYTHONPATH=$PWD
timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > gpurun_out/bench_r02i.json 2> gpurun_out/bench_r02i.err
python -c "
import json; d=json.load(open('gpurun_out/bench_r02i.json'))
print('C2 value %.4g ms/step %.1f frac %.3f' % (d['value'], d['ms_per_step'], d['roofline']['frac']))
for k,v in d['config']['per_query'].items(): print('  %-16s %9.2f ms' % (k, v['time_to_count_ms']))
"
timeout 600 python scripts/configs_probe.py 4 prism 64 0 0 10 0 stats > gpurun_out/diag_c4.log 2>&1; cat gpurun_out/diag_c4.log
for b in 3 4 5; do
  timeout 1500 python bench.py --config $b --steps 1 --warmup 1 --no-e2e --cpu-sample-world 200001 > gpurun_out/bench_r02i_c$b.json 2> gpurun_out/bench_r02i_c$b.err
  python -c "
import json; d=json.load(open('gpurun_out/bench_r02i_c$b.json'))
print('C$b value %.4g ms/step %.1f frac %.3f' % (d['value'], d['ms_per_step'], d['roofline']['frac']))
for k,v in d['config']['per_query'].items(): print('  %-16s %9.2f ms  count %d  tail(first/mean/last ms) %s' % (k, v['time_to_count_ms'], v['count'], v['warp_exit_ms_first_mean_last_stats_run']))
" || tail -5 gpurun_out/bench_r02i_c$b.err
done
