#!/bin/bash
# run arbitrary commands (one per argument) after the build; outputs cmd_<i>.log
TAG=${1:-cmd}
OUT=gpurun_out/$TAG
mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
shift
i=0
for c in "$@"; do
  i=$((i+1))
  echo "$i: $c" >> $OUT/configs.txt
  timeout 900 bash -c "$c" > $OUT/cmd_$i.log 2>&1
  echo "exit $?" >> $OUT/cmd_$i.log
done
echo done > $OUT/DONE
