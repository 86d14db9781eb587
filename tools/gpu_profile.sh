#!/bin/bash
# ncu captures of the round (profile_round.sh), summarised ON the box (the
# .ncu-rep files exceed what gpurun copies back): summaries and the launch list
# land in gpurun_out/prof_summary/, the raw reports are deleted except the
# cold-cache SpMV / ring captures' raw pages (already in the summary).
mkdir -p gpurun_out/prof_summary
bash tools/profile_round.sh ${1:-hpccg256}
PROFILES_OUT=gpurun_out/prof_summary python tools/summarize_profiles.py ${TAG:-r2} ${1:-hpccg256} > gpurun_out/prof_summary/summary.txt 2>&1
for r in gpurun_out/*.ncu-rep; do
  ncu -i "$r" --page details --csv > "gpurun_out/prof_summary/$(basename $r .ncu-rep)_details.csv" 2>/dev/null
done
rm -f gpurun_out/*.ncu-rep
du -sh gpurun_out
