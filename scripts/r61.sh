# round 2: compute-sanitizer memcheck / racecheck / synccheck over the small GPU parity cases
bash scripts/sanitize.sh
