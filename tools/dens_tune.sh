# A/B of the density kernel's shape knobs on C2 (points per plane, planes per CTA, y chunks)
for cfg in "18 1 1" "36 1 1" "18 2 1" "36 2 1" "12 5 1" "12 5 2" "8 5 2" "18 2 2" "24 2 1" "9 5 2" "12 2 1" "8 7 2"; do
 set -- $cfg
 LFD_DENS_PX=$2 LFD_DENS_YC=$3 python tools/tune.py --knob LFD_DENS_ZCMAX --values $1 --steps 20 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('zc', d['value'], 'px', $2, 'yc', $3, d['ms_per_launch'].get('density'))
"
done
