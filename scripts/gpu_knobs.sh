mkdir -p gpurun_out
run() { env "$@" timeout 300 python bench.py --no-corun --no-c4 --no-plans --no-fusion --no-cpu-baseline --no-e2e --steps 200 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('$*', round(d['ms_per_step']*1e3,2), round(d['roofline']['eager']['kernel_ms']*1e3,2))"; }
for rep in 1 2; do
for k in ${KNOBS:-X=0}; do run $k; done
done
