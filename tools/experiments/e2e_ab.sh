for r in 1 2; do for v in ring_off ring_on; do
  CGCM_LIBDIR=$PWD/build/ab/$v timeout 300 python bench.py --no-cpu-baseline --steps 3 > gpurun_out/e2e_$v.log 2>&1
  python -c "import json,sys; d=json.loads([l for l in open('gpurun_out/e2e_$v.log') if l.startswith('{')][-1]); print('$v', d['roofline']['fwd_ms_per_launch'], d['e2e']['ms_per_step'], d['clocks'])"
  CGCM_LIBDIR=$PWD/build/ab/$v timeout 300 python tools/bench_configs.py B 2>&1 | cut -c1-80
done; done
