python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in "18 1 1" "18 1 2" "9 1 1" "9 1 2" "12 1 1" "24 1 1" "36 1 1" "18 2 1"; do
 set -- $cfg
 LFD_DENS_ZCMAX=$1 LFD_DENS_PX=$2 LFD_DENS_YC=$3 timeout 300 python bench.py --no-cpu-baseline --no-e2e --no-sc --no-sp --steps 50 2>/dev/null > gpurun_out/dab.json
 python -c "
import json; d=json.load(open('gpurun_out/dab.json')); print('zc $1 px $2 yc $3 density', round(d['kernels']['density']['ms_per_launch'],4), 'step', round(d['ms_per_step'],4))"
done
