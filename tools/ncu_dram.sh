#!/bin/bash
# DRAM bytes + duration of every probe-family launch of one bench run:
#   bash tools/ncu_dram.sh <tag> <workload> [bench args...]
T=$1; W=$2; shift 2
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct --clock-control none \
    -k regex:"k_probe|k_deferred|k_fixup|k_move|k_pp|k_multi" -c 12 --csv --log-file gpurun_out/${T}_dram_${W}.csv \
    python bench.py --workload $W --profile --steps 2 --warmup 1 "$@" > /dev/null 2>&1
python - gpurun_out/${T}_dram_${W}.csv <<'PY'
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
i = next(k for k, r in enumerate(rows) if r and r[0] == "ID")
hdr = rows[i]; d = collections.OrderedDict()
for r in rows[i + 1:]:
    x = dict(zip(hdr, r)); d.setdefault((x["ID"], x["Kernel Name"][:40]), {})[x["Metric Name"]] = x["Metric Value"]
for k, v in d.items(): print(k, v)
PY
