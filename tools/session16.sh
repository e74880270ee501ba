set -u
for seg in 1 0 1 0; do
GRANII_GATBWD_SEG=$seg CASES="17:100:256;16:256:47" TUNES="def" timeout 900 python tools/gatbwd_sweep.py products 2>&1 | tail -2 | sed "s/^/seg=$seg /"
done
