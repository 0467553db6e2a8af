#!/bin/bash
# On the GPU box: Table 5 / Fig 5 analogue — per breakdown variant (Fig 6) of the Box-2D9P pass
# kernel, the shared-memory bank conflicts, shared wavefronts, global sectors per request
# (coalescing) and DRAM bytes of one main-pass launch (ncu, cold cache, serialised).
OUT=gpurun_out/breakdown_ncu.csv
NCU=/usr/local/cuda/bin/ncu
M=gpu__time_duration.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum,l1tex__t_requests_pipe_lsu_mem_global_op_st.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active
: > $OUT
B="python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-comparator"
run() {  # tag kernel-regex skip args...
  local tag=$1 kre=$2 skip=$3; shift 3
  $NCU --metrics $M --clock-control none -k regex:$kre -s $skip -c 1 --csv $B "$@" 2>/dev/null | \
    sed -n '/"ID"/,$p' | sed "s/^/\"$tag\",/" >> $OUT
}
run direct k_direct2d 3 --engine direct
run I k_s2r_explicit_fma 3 --engine tc_s2r --s2r-variant I
run I_transform k_s2r_explicit_transform 3 --engine tc_s2r --s2r-variant I
for v in II III IV V; do run $v k_s2r2d 3 --engine tc_s2r --s2r-variant $v; done
run tc_tile k_tile2d 3
python - <<'PY'
import csv, collections
rows = list(csv.reader(open("gpurun_out/breakdown_ncu.csv")))
d = collections.OrderedDict()
for r in rows:
    if len(r) < 5 or r[1] == "ID":
        continue
    tag, name, unit, val = r[0], r[-3], r[-2], r[-1]
    d.setdefault(tag, {})[name] = (val, unit)
for tag, m in d.items():
    print(tag, {k.split("__")[1][:40]: v[0] for k, v in m.items()})
PY
