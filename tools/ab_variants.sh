for i in 1 2; do
for L in "" paper_conf_ipps_lizzh12_b200/libstarsim_OLD.so; do
STARSIM_LIB=$L timeout 300 python bench.py --steps 20 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); v=d['variants']; print('$L', round(d['ms_per_step']*1e3,1), round(v['atomic']['ms_per_step']*1e3,1), round(v['lut']['ms_per_step']*1e3,1), round(v.get('atomic_circle',{}).get('ms_per_step',0)*1e3,1))"
done; done
