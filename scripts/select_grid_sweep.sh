for C in 3 2; do for G in 74 148 296 592; do
  LOWDIFF_SELECT_GRID=$G timeout 300 python bench.py --config $C --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/selg_${C}_$G.json 2>/dev/null
  python -c "
import json;d=json.load(open('gpurun_out/selg_${C}_$G.json'))
print('C$C grid $G', round(d['kernels']['compress_select']['ms_per_step']/d['kernels']['compress_select']['launches_per_step']*1e3,1), 'us/launch')"
done; done
