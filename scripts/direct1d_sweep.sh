for V in 4 8 16; do for PF in 0 1; do
 CSX_DIRECT1D_V=$V CSX_DIRECT1D_PF=$PF timeout 300 python -m pytest tests -m gpu -q -k "direct" 2>&1 | tail -1 | sed "s/^/tests V=$V PF=$PF: /"
done; done > gpurun_out/d1_tests.log
for cfg in heat1d_10240000 1d5p_10240000; do
 for V in 4 8 16; do for PF in 0 1; do for F in 0 6; do
   FA=""; [ $F -gt 0 ] && FA="--fuse $F"
   echo "cfg=$cfg V=$V PF=$PF F=$F $(CSX_DIRECT1D_V=$V CSX_DIRECT1D_PF=$PF timeout 120 python bench.py --config $cfg --engine direct $FA --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-comparator 2>&1 | tail -1 | python -c 'import sys,json; d=json.loads(sys.stdin.read()); print(round(d["value"],1), d["config"].get("fuse_steps"))' 2>&1 | tail -1)"
 done; done; done
done > gpurun_out/d1_sweep.txt 2>&1
cat gpurun_out/d1_tests.log gpurun_out/d1_sweep.txt
