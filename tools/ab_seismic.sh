for rep in 1 2; do for spec in "default" "default+SAFARA_SEISMIC_LDG=1"; do
lib=${spec%%+*}; env=${spec#*+}; [ "$env" = "$spec" ] && env=""
if [ "$lib" = "default" ]; then L=""; else L="SAFARA_LIB=ablibs/$lib.so"; fi
env $L $env timeout 200 python bench.py --workload seismic_dz --steps 100 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print('$spec', round(d['ms_per_step']*1e3,2), 'us', round(d['roofline']['frac'],3), d['clocks']['sm_mhz'])"
done; done
