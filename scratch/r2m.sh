cd $GRAFT_REPO_ROOT
N="timeout 600 ncu --set full --import-source on --clock-control none --kernel-name-base demangled"
$N -k "regex:acs::k_esc<" -s 1 -c 1 -o gpurun_out/r2m_esc_cfg3_f64 python scratch/one.py cfg3 f64 > gpurun_out/r2m_p1.log 2>&1
$N -k "regex:acs::k_esc<" -s 1 -c 1 -o gpurun_out/r2m_esc_cfg5_f64 python scratch/one.py cfg5 f64 > gpurun_out/r2m_p2.log 2>&1
timeout 600 python tools/table3.py > gpurun_out/r2m_table3.md 2> gpurun_out/r2m_table3.err
