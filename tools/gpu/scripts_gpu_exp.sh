#!/bin/bash
# experiment session: run the commands in exp_cmds.txt (one per line) with logs under gpurun_out/exp/
cd "$GRAFT_REPO_ROOT" || exit 1
mkdir -p gpurun_out/exp
i=0
while IFS= read -r cmd; do
  [ -z "$cmd" ] && continue
  i=$((i+1))
  echo "### $cmd" > gpurun_out/exp/$i.log
  timeout 900 bash -c "$cmd" >> gpurun_out/exp/$i.log 2>&1
  echo "rc=$?" >> gpurun_out/exp/$i.log
done < exp_cmds.txt
echo done
