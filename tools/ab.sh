#!/bin/bash
# Same-box A/B: tools/ab.sh SPEC [SPEC ...] -- times tools/quick.py (or $SCRIPT)
# for each SPEC = <lib.so>[:VAR=VAL[,VAR=VAL...]] (env knobs of libsat),
# interleaved twice so that pool-to-pool box variation cancels.
for rep in $(seq 1 ${REPS:-2}); do
  for SPEC in "$@"; do
    L=${SPEC%%:*}
    ENVS=""
    [[ "$SPEC" == *:* ]] && ENVS=${SPEC#*:}
    echo "== $L${ENVS:+[$ENVS]} (rep $rep)"
    env ${ENVS//,/ } SAT_LIBRARY=$L timeout 300 python ${SCRIPT:-tools/quick.py} ${STEPS:-10}
  done
done
