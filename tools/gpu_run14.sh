for c in tunnel4 sphere3 sphere_tab1_s3 cavity4_kbc; do
  for v in paper volumetric; do
    timeout 400 python bench.py --config $c --variant $v --steps 30 --no-cpu-baseline > gpurun_out/r01v_${c}_${v}.json 2> gpurun_out/r01v_${c}_${v}.err
  done
done
python tools/sweep_table.py gpurun_out/r01v_*.json
tail -3 gpurun_out/r01v_tunnel4_volumetric.err
