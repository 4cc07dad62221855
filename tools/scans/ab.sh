# same-box A/B: tools/scans/ab.sh "<shapes>" PAIR lib1 lib2 ...
L=paper_conf_cluster_chenwttm18_b200
S="$1"; PAIR=$2; shift 2
for rep in 1 2; do for v in "$@"; do
echo "== $v rep $rep"; SAT_LIBRARY=$L/$v.so python tools/shape_scan.py $PAIR $S
done; done
