# A/B of seismic dz variants (bench.py --workload seismic_dz, 256^3); args: SPEC ... (LIB[+ENV=V])
for rep in 1 2 3; do for spec in "$@"; do
lib=${spec%%+*}; env=${spec#*+}; [ "$env" = "$spec" ] && env=""
if [ "$lib" = "default" ]; then L=""; else L="SAFARA_LIB=ablibs/$lib.so"; fi
env $L $env timeout 200 python bench.py --workload seismic_dz --steps 100 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print('$spec', round(d['ms_per_step']*1e3,2), 'us', round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['clocks'].get('power_w_max'))"
done; done
