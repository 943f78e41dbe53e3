#!/bin/bash
# SASS evidence for the copy kernels (no GPU needed): resource usage (registers, spills =
# LOCAL / STACK), instruction-class counts, and excerpts around the bulk-copy instructions.
# Usage: scripts/sass_evidence.sh > profiles/r02/sass_copy_kernels.txt
set -e
LIB=${1:-paper_conf_isca_fenghzly025_b200/libwind_kv.so}
echo "# cuobjdump of $LIB ($(cuobjdump --version | tail -1))"
echo "# built by __graft_entry__.build(): nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo"
echo
echo "## resource usage (REG = registers/thread; STACK / LOCAL = spill space: 0 = no spills)"
cuobjdump --dump-resource-usage "$LIB" | grep -A1 -E "Function .*(tma_copy|simt_copy|flag_bump)" | sed 's/^ *//'
TMP=$(mktemp)
cuobjdump -sass "$LIB" > "$TMP"
PAT='\b(UBLKCP[A-Z.0-9]*|UTMA[A-Z.0-9]*|SYNCS\.[A-Z.0-9]+|FENCE\.[A-Z.]+|MEMBAR\.[A-Z.]+|REDG[A-Z.0-9]*|ATOMG\.[A-Z.0-9]+|VOTE\.[A-Z]+|POPC|SHFL\.[A-Z]+|LDG\.[A-Z.0-9]+|STG\.[A-Z.0-9]+|NANOSLEEP|ACQBULK|DEPBAR[A-Z.0-9]*|CCTL[A-Z.]*|STL[A-Z.0-9]*|LDL[A-Z.0-9]*)\b'
for k in tma_copy_kernel simt_copy_kernel; do
  echo
  echo "## $k: instruction classes (count)"
  awk -v k="$k" '/Function :/{on = index($0, k) > 0} on' "$TMP" > "$TMP.$k"
  grep -oE "$PAT" "$TMP.$k" | sort | uniq -c | sort -rn
  echo "## $k: total SASS lines $(grep -cE '^ +/\*[0-9a-f]{4}\*/' "$TMP.$k"); local-memory (spill) instructions: $(grep -cE '\b(STL|LDL)\b' "$TMP.$k" || true)"
done
echo
echo "## tma_copy_kernel: excerpts (bulk global->shared load with mbarrier complete_tx, shared->global store, bulk-group wait)"
grep -nE "UBLKCP|SYNCS|DEPBAR" "$TMP.tma_copy_kernel" | head -40 | sed 's/ *\/\* 0x[0-9a-f]* \*\///'
echo
echo "## simt_copy_kernel: excerpts (16-B vector loads / stores)"
grep -nE "LDG.E.NA.128|STG.E.NA.128" "$TMP.simt_copy_kernel" | head -16 | sed 's/ *\/\* 0x[0-9a-f]* \*\///'
rm -f "$TMP" "$TMP".*
