CONFIGS="m1 m2 m3" bash tools/ab_k1b.sh base warpred=FFSVA_K1_WARPRED=1 > gpurun_out/ab_k1c.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sdd -s 40 -c 1 -o gpurun_out/prof_k1_m2_refpre -f \
    python bench.py --config m2 --steps 20 --warmup 3 --no-e2e --no-cpu-baseline --online "" --online-tyolo "" > gpurun_out/ncu_k1c.log 2>&1
echo "ncu rc=$?" >> gpurun_out/ab_k1c.log
