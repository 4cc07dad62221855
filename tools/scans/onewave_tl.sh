# Where does a one-wave 8u image (8192^2) spend its time?  Timeline + look-back profile, CL 4 and 8.
L=paper_conf_cluster_chenwttm18_b200
for cl in 4 8; do
  rm -f gpurun_out/tl_ow_$cl.txt
  STEPS=1 SAT_CLUSTER=$cl SAT_TIMELINE_OUT=gpurun_out/tl_ow_$cl.txt SAT_LIBRARY=$L/libsat_tl.so timeout 60 python tools/shape_scan.py 0 8192x8192
  python tools/tl_analyze.py gpurun_out/tl_ow_$cl.txt
  echo "== prof CL=$cl"; STEPS=2 SAT_CLUSTER=$cl SAT_LIBRARY=$L/libsat_prof.so timeout 60 python tools/shape_scan.py 0 8192x8192 2>&1 | tail -6
done
