set -u
for v in new old new old; do
  if [ $v = old ]; then D=tmp_ab; else D=.; fi
  CASES="17:100:256;16:256:47" TUNES="def" timeout 900 python $D/tools/gatbwd_sweep.py products 2>&1 | tail -2 | sed "s/^/$v /"
done
