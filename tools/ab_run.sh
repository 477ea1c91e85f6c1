#!/bin/bash
# A/B of libspade.so builds: LIBS="a.so b.so" WLS="c3 c4" REPS=2 bash tools/ab_run.sh [extra bench args]
# (restores the in-tree library afterwards)
cp paper_conf_icde_doraiswamyf22_b200/libspade.so /tmp/libspade_orig.so
for r in $(seq ${REPS:-1}); do
for L in $LIBS; do
  cp "$L" paper_conf_icde_doraiswamyf22_b200/libspade.so
  for wl in ${WLS:-c3}; do
    timeout 600 python bench.py --workload $wl --no-e2e --no-cpu-baseline --no-parity --steps ${STEPS:-20} --warmup 3 "$@" > /tmp/ab_$wl.json 2>/tmp/ab_$wl.err \
    && python -c "import json; d=json.load(open('/tmp/ab_$wl.json')); r=d['roofline']; st=d.get('stages_ms') or {}; print('$(basename $L)', '$wl', 'kernel %.3f ms' % r['kernel_ms'], 'step %.3f ms' % d['ms_per_step'], 'frac %.3f' % r['frac'], ' '.join('%s=%.2f' % (k[:6], v) for k, v in st.items()), d['check'])" \
    || { echo "$(basename $L) $wl FAILED"; tail -3 /tmp/ab_$wl.err; }
  done
done
done
cp /tmp/libspade_orig.so paper_conf_icde_doraiswamyf22_b200/libspade.so
