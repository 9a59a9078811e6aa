for c in sphere_tab1_s1 sphere_tab1_s2 sphere_tab1_s3 tunnel4; do
  p=fp64; [ $c = tunnel4 ] && p=fp32
  for s in fig4b fig4c fig4d fig4e fig4f unfused cta_gather fused; do
    timeout 300 python bench.py --config $c --precision $p --schedule $s --steps 20 --no-cpu-baseline --no-secondary --no-ncu-traffic > gpurun_out/r02c_fig9_${c}_${s}.json 2>/dev/null
  done
done
python tools/ablation_table.py gpurun_out/r02c_fig9 > gpurun_out/r02c_fig9_ablation.txt
cat gpurun_out/r02c_fig9_ablation.txt
