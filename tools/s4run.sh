# correctness of nk2_select4 / nk3_merge4 in isolation (tools/sort4_check.cu)
for a in "200000 26112 0" "200000 26112 1" "200000 26112 2" "1000003 26112 3" "4194304 26112 0" "16777216 1671168 0" "16777216 3342336 1" "9000001 26112 2" "9000001 417792 1"; do
  echo "== $a"; timeout 60 ./tools/sort4_check $a 2>&1 | grep -E "mismatch|stall|error" | head -4
  echo "-- exact"; timeout 60 ./tools/sort4_check_exact $a 2>&1 | grep -E "mismatch|stall|error" | head -4
done
