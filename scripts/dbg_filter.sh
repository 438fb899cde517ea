for cfg in "" "GCSM_NO_FILTER3=1" "GCSM_NO_HOIST=1" "GCSM_NO_FILTER3=1 GCSM_NO_HOIST=1"; do
  echo "== $cfg" >> gpurun_out/dbg.txt
  env $cfg python -m pytest tests -m gpu -q -k "six_vertex_queries or symmetry_breaking_on_off or motif_census" 2>&1 | tail -4 >> gpurun_out/dbg.txt
done
