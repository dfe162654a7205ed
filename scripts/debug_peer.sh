for args in "2 9000 uniform 1 0" "2 9000 uniform 0 0" "2 9000 plummer 1 0" "4 30001 plummer 0 0" "2 9000 uniform 1 1" "2 20000 disks 1 0"; do
  timeout 60 python scripts/debug_peer.py $args 2>&1 | tail -1
done
