O=gpurun_out/prof; R=/tmp/prof_reps
mkdir -p $O
if [ ! -f $R/p4_16384x16384x1.ncu-rep ]; then bash tools/scans/profile_final.sh; exit; fi
cp -r profiles/. /tmp/keep_profiles 2>/dev/null
python tools/ncu_summary.py r01 $R/*.ncu-rep --launches gpurun_out/launches_prev.csv > $O/summary.log 2>&1
cp profiles/r01_ncu.md profiles/ncu_summary.json $O/
