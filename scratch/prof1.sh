set -x
cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" || exit 1
N="ncu --set full --import-source on --clock-control none"
$N -k regex:k_dict -s 1 -c 1 -o gpurun_out/r2a_dict_cfg2_f64 python scratch/one.py cfg2 f64 dict > gpurun_out/r2a_p1.log 2>&1
$N -k regex:k_hash -s 1 -c 1 -o gpurun_out/r2a_hash_cfg2_f64 python scratch/one.py cfg2 f64 > gpurun_out/r2a_p2.log 2>&1
$N -k regex:k_esc -s 1 -c 1 -o gpurun_out/r2a_esc_cfg3_f64 python scratch/one.py cfg3 f64 > gpurun_out/r2a_p3.log 2>&1
$N -k regex:k_esc -s 1 -c 1 -o gpurun_out/r2a_esc_cfg5_f64 python scratch/one.py cfg5 f64 > gpurun_out/r2a_p4.log 2>&1
ls -la gpurun_out
