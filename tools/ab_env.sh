#!/bin/bash
# A/B of library env switches on one probe:  tools/ab_env.sh OUT "ENV1" "ENV2" ... -- probe args
# each ENV string is a space-separated list of VAR=VALUE (or "-" for none)
out=$1; shift
envs=()
while [ "$1" != "--" ]; do envs+=("$1"); shift; done
shift
for e in "${envs[@]}"; do
  echo "### env: $e" >> "$out"
  if [ "$e" = "-" ]; then python "$@" >> "$out" 2>&1; else env $e python "$@" >> "$out" 2>&1; fi
done
