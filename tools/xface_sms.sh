#!/bin/bash
# C4 x-face pack/unpack by SM cap and kernel family (register word table vs cp.async staging)
for sms in 16 32 148; do for k in 2 4; do
  echo "sms=$sms kind=$k $(DT_MAX_SMS=$sms DT_FORCE_KERNEL=$k timeout 120 python tools/kbench.py --configs C4x --reps 10 2>&1 | tail -1)"
done; done
